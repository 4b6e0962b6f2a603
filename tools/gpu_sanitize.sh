#!/bin/bash
# compute-sanitizer memcheck / synccheck / racecheck over every kernel variant (tools/sanitize_run.py)
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for tool in memcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py > gpurun_out/r03_sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/r03_sanitize_$tool.log
done
