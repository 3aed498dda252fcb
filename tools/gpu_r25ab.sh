for rep in 1 2; do for v in old new; do
SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 900 python bench.py --workload rmat25 --hybrid 2 --steps 30 --warmup 3 --no-cpu-baseline --no-variants --spmm "" > gpurun_out/r25_$v.json 2>gpurun_out/r25_$v.err
python -c "import json; d=json.load(open('gpurun_out/r25_$v.json')); print('$v', round(d['roofline']['kernel_ms'],3), 'cusparse', round(d['cusparse_csr']['ms'],3))"
done; done
