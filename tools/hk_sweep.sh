for cfg in ${HK_CFGS:-"128 2" "256 1"}; do
  set -- $cfg
  echo "NN=$1 T=$2" >> gpurun_out/hk8s.log
  POLYCONV_HK_NN=$1 POLYCONV_HK_T=$2 HK_DBGS="0" timeout 120 python tools/hk_trace.py 256 256 14 14 256 3 3 >> gpurun_out/hk8s.log 2>&1
  POLYCONV_HK_NN=$1 POLYCONV_HK_T=$2 HK_DBGS="0" timeout 120 python tools/hk_trace.py 256 512 7 7 512 3 3 >> gpurun_out/hk8s.log 2>&1
  POLYCONV_HK_NN=$1 POLYCONV_HK_T=$2 HK_DBGS="0" timeout 120 python tools/hk_trace.py 32 128 28 28 128 3 3 >> gpurun_out/hk8s.log 2>&1
  POLYCONV_HK_NN=$1 POLYCONV_HK_T=$2 HK_DBGS="0" timeout 120 python tools/hk_trace.py 256 128 28 28 128 3 3 >> gpurun_out/hk8s.log 2>&1
done
