#!/bin/bash
# Round-2 ncu evidence: full captures of mac_hankel at the bench shape (conv3_x N=32) and the four
# gate layers (ResNet-50 N=256 stride-1 3x3), a stride-2 layer (phase mode), the stem, the FFT solver's
# kernels at ResNet-50 l4 (FP32, NCU_FFT=1), and
# the launch list of a short bench run.  Usage (GPU box, repo root): bash tools/gpu_ncu_r02.sh
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
run() {  # name, kernel regex, command...
  local name=$1 rx=$2; shift 2
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:$rx -s 2 -c 1 -o gpurun_out/r02_$name "$@" > gpurun_out/r02_$name.log 2>&1
  echo "$name rc=$?"
}
run hk_conv3x mac_hankel python tools/hk_one.py 32 128 28 28 128 3 3
run hk_l1 mac_hankel python tools/hk_one.py 256 64 56 56 64 3 3
run hk_l2 mac_hankel python tools/hk_one.py 256 128 28 28 128 3 3
run hk_l3 mac_hankel python tools/hk_one.py 256 256 14 14 256 3 3
run hk_l4 mac_hankel python tools/hk_one.py 256 512 7 7 512 3 3
run hk_l3s2 mac_hankel python tools/hk_one.py 256 256 28 28 256 3 3 2 1
run hk_stem mac_hankel python tools/hk_one.py 256 3 224 224 64 7 7 2 3
if [ "${NCU_FFT:-0}" = 1 ]; then
  for k in fft_rows_fwd fft_filter_eval fft_contract fft_rows_inv; do
    run fft_l4_$k $k python tools/fft_one.py 256 512 7 7 512 3 3
  done
fi
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_bench.csv \
  python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cudnn --no-gate --no-by-math > gpurun_out/r02_launches_bench.log 2>&1
echo "launches rc=$?"
