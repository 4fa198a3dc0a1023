#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on smoke() and tools/sanitize_paths.py
#   gpurun --timeout 2400 -- 'bash tools/sanitize.sh'   (logs in gpurun_out/san_*.log)
set -u
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/san_smoke_$tool.log 2>&1
  echo "smoke $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san_smoke_$tool.log)"
  timeout 900 compute-sanitizer --tool $tool python tools/sanitize_paths.py > gpurun_out/san_paths_$tool.log 2>&1
  echo "paths $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san_paths_$tool.log)"
done
