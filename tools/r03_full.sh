# full GPU suite + smoke + bench (all records) + ResNet-50 stack + layer sweeps + ncu launch list of the bench
set -u
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r03_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03_smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/r03_smoke.log
timeout 900 python bench.py > gpurun_out/r03_bench.json 2> gpurun_out/r03_bench.err; echo "bench rc=$?"; tail -c 300 gpurun_out/r03_bench.json
timeout 600 python bench.py --workload resnet50 --no-cpu-baseline > gpurun_out/r03_bench_resnet50.json 2>> gpurun_out/r03_bench.err; echo "bench r50 rc=$?"
timeout 900 python tools/layer_sweep.py resnet50 > gpurun_out/r03_sweep_resnet50_n256.jsonl 2>&1; echo "sweep r50 rc=$?"
timeout 900 python tools/layer_sweep.py vgg16 > gpurun_out/r03_sweep_vgg16_n64.jsonl 2>&1; echo "sweep vgg rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r03_launches_bench.csv \
  python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cudnn --no-gate --no-by-math > gpurun_out/r03_launches_bench.log 2>&1; echo "launches rc=$?"
