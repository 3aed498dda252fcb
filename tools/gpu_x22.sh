for c in 0 2097152 1048576; do
  if [ $c = 0 ]; then unset SPADEN_XSEG_COLS; else export SPADEN_XSEG_COLS=$c; fi
  timeout 600 python bench.py --workload rmat22 --hybrid 3 --steps 200 --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['config']['residual_parts'], round(d['roofline']['kernel_ms'],4))"
done
