# full GPU suite + smoke + bench (all records) + ResNet-50 stack + layer sweeps + ncu launch list + ncu full captures
set -u
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r03_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03_smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/r03_smoke.log
timeout 900 python bench.py > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err; echo "bench rc=$?"
timeout 600 python bench.py --workload resnet50 --no-cpu-baseline > gpurun_out/r03_bench_resnet50.json 2>> gpurun_out/r03_bench.err; echo "bench r50 rc=$?"
timeout 900 python tools/layer_sweep.py resnet50 > gpurun_out/r03_sweep_resnet50_n256.jsonl 2>&1; echo "sweep r50 rc=$?"
timeout 900 python tools/layer_sweep.py vgg16 > gpurun_out/r03_sweep_vgg16_n64.jsonl 2>&1; echo "sweep vgg rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r03_launches_bench.csv \
  python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cudnn --no-gate --no-by-math > gpurun_out/r03_launches_bench.log 2>&1; echo "launches rc=$?"
run() { local name=$1 rx=$2; shift 2
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:$rx -s 2 -c 1 -o gpurun_out/r03_$name "$@" > gpurun_out/r03_$name.log 2>&1; echo "$name rc=$?"; }
run hk_conv3x mac_hankel python tools/hk_one.py 32 128 28 28 128 3 3
run hk_l4 mac_hankel python tools/hk_one.py 256 512 7 7 512 3 3
run hk_l1 mac_hankel python tools/hk_one.py 256 64 56 56 64 3 3
run hk_stem mac_hankel python tools/hk_one.py 256 3 224 224 64 7 7 2 3


run 1x1_l4x mac_1x1 python tools/hk_one.py 256 512 7 7 2048 1 1 1 0
