# FP32 direct kernel: GPU tests, bench conv3x FP32, per-layer FP32 comparison vs FFT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r03_pytest_gpu.log
timeout 600 python bench.py --math fp32 --no-cpu-baseline --no-gate --no-by-math --steps 50 > gpurun_out/r03_bench_fp32.json 2> gpurun_out/r03_bench_fp32.err; echo "bench rc=$?"
timeout 900 python tools/fp32_cmp.py ${CMP:-all} > gpurun_out/r03_fp32_cmp.jsonl 2>&1; echo "cmp rc=$?"
