#!/bin/bash
# GPU test suite (+ smoke), logs under gpurun_out/tests
mkdir -p gpurun_out/tests
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/tests/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/tests/smoke.log
timeout ${T:-1800} python -m pytest tests -m gpu -q -x ${K:+-k "$K"} --timeout 900 > gpurun_out/tests/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/tests/pytest_gpu.log
tail -5 gpurun_out/tests/pytest_gpu.log; tail -2 gpurun_out/tests/smoke.log
