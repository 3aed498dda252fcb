#!/bin/bash
# compute-sanitizer (memcheck / racecheck / synccheck / initcheck) over tools/sanitize_run.py
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --target-processes all python tools/sanitize_run.py > gpurun_out/sanitizer_$tool.log 2>&1; echo "rc=$?" >> gpurun_out/sanitizer_$tool.log
done
for tool in memcheck racecheck synccheck initcheck; do echo "== $tool"; tail -4 gpurun_out/sanitizer_$tool.log; done
