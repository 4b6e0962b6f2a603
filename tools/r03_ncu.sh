# source-level ncu captures of mac_hankel at l2 and l3 (where do the loaders / epilogue stall)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for L in "l2 256 128 28 28 128 3 3" "l3 256 256 14 14 256 3 3"; do
  set -- $L; name=$1; shift
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:mac_hankel -s 2 -c 1 -o gpurun_out/r03_hk_$name python tools/hk_one.py "$@" > gpurun_out/r03_hk_$name.log 2>&1
  echo "$name rc=$?"
done
