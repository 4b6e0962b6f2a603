python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
for C in 8 16 32; do
  POLYCONV_F32_CC=$C timeout 600 python tools/fp32_cmp.py resnet50 > gpurun_out/r03_fp32cc_$C.jsonl 2>&1
done
