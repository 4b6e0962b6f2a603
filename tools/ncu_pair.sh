python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mac_pair -s 3 -c 1 -o gpurun_out/${1:-pair} \
    python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-cudnn > gpurun_out/${1:-pair}_ncu.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/${1:-pair}_ncu.log
