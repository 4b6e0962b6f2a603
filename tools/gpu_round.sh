#!/bin/bash
# One gpurun session: build, GPU tests, bench, ncu launch list + full capture of the MAC.
# Usage (from the repo root on the GPU box): bash tools/gpu_round.sh [tests|bench|ncu|all] [tag]
set -u
what=${1:-all}; tag=${2:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${tag}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${tag}_build.log 2>&1 || { tail -30 gpurun_out/${tag}_build.log; exit 1; }
if [[ $what == tests || $what == all ]]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${tag}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/${tag}_pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1; echo "smoke rc=$?"; tail -4 gpurun_out/${tag}_smoke.log
fi
if [[ $what == bench || $what == all ]]; then
  timeout 600 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?"; cat gpurun_out/${tag}_bench.json; tail -3 gpurun_out/${tag}_bench.err
  for m in tf32 fp32; do
    timeout 600 python bench.py --math $m --no-cpu-baseline > gpurun_out/${tag}_bench_$m.json 2>> gpurun_out/${tag}_bench.err; echo "bench $m rc=$?"
  done
fi
if [[ $what == ncu || $what == all ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cudnn > gpurun_out/${tag}_ncu_bench.log 2>&1; echo "ncu launches rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:mac_pair -s 3 -c 1 -o gpurun_out/${tag}_mac_pair \
    python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-cudnn > gpurun_out/${tag}_ncu_full.log 2>&1; echo "ncu full rc=$?"
  timeout 600 ncu --set full --clock-control none -k regex:pack -s 3 -c 1 -o gpurun_out/${tag}_pack \
    python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-cudnn > gpurun_out/${tag}_ncu_pack.log 2>&1; echo "ncu pack rc=$?"
fi
