#!/bin/bash
# health check at HEAD: smoke, pytest -m gpu, default bench lines (fp32 / fp16)
O=gpurun_out/chk; mkdir -p $O
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_fp32.json 2> $O/bench_fp32.err
timeout 600 python bench.py --dtype fp16 --spmm "" --spmm-tc "" --no-cpu-baseline > $O/bench_fp16.json 2> $O/bench_fp16.err
tail -3 $O/pytest_gpu.log; tail -2 $O/smoke.log
python - <<'PY'
import json
for f in ['gpurun_out/chk/bench_fp32.json', 'gpurun_out/chk/bench_fp16.json']:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, d['value'], d['roofline']['frac'], d.get('convert'))
    except Exception as e:
        print(f, 'ERR', e)
PY
