python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python tools/kernel_cmp.py resnet50 8 > gpurun_out/r03_kcmp_resnet50.jsonl 2>&1; echo "kcmp rc=$?"
timeout 900 python tools/kernel_cmp.py sweep 6 > gpurun_out/r03_kcmp_sweep.jsonl 2>&1; echo "kcmp sweep rc=$?"
timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > gpurun_out/r03_bench_resnet50.json 2>/dev/null; echo "r50 rc=$?"
