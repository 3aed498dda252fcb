#!/bin/bash
# default bench line (+clocks), fp16 line, reference arm; logs under gpurun_out/bench
mkdir -p gpurun_out/bench
timeout 900 python bench.py ${ARGS} > gpurun_out/bench/default.json 2> gpurun_out/bench/default.err
timeout 900 python bench.py --dtype fp16 --spmm "" ${ARGS} > gpurun_out/bench/fp16.json 2> gpurun_out/bench/fp16.err
timeout 600 python bench.py --impl reference > gpurun_out/bench/reference.json 2> gpurun_out/bench/reference.err
python - <<'PY'
import json
for f in ("default", "fp16", "reference"):
    try:
        d = json.load(open(f"gpurun_out/bench/{f}.json"))
        print(f, round(d["value"], 1), d.get("roofline", {}).get("frac"), d.get("cusparse_csr", {}) and {k: v for k, v in d["cusparse_csr"].items() if k in ("ms", "best", "speedup_spaden_vs_cusparse")}, d.get("cpu_baseline", {}) and (d["cpu_baseline"]["value"], d["cpu_baseline"]["cores"]), d.get("convert"), d.get("e2e", {}).get("value"))
    except Exception as e:
        print(f, "ERR", e)
PY
