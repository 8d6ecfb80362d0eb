set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "table" > gpurun_out/pytest_r02t2.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_r02t2.log
for rep in 1 2; do
for v in new old; do
  if [ $v = old ]; then export OLAP_LIB=abv/oldtable.so; else unset OLAP_LIB; fi
  timeout 300 python bench.py --workload T --no-cpu-baseline --e2e-steps 0 > gpurun_out/ab_r02t2_${v}_$rep.log 2>&1
  tail -1 gpurun_out/ab_r02t2_${v}_$rep.log > gpurun_out/ab_r02t2_${v}_$rep.jsonl
done
done
unset OLAP_LIB
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
    -k regex:table_scan --csv --log-file gpurun_out/traffic_r02t2_T.csv \
    python bench.py --workload T --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
echo done
