# Session-4: queries scanned in op-grouped order (table_order_kernel).
# Table parity, then an A/B of T against abvar/head.so (the previous table.cu), alternating.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4e.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "table or tpcds or smoke" > gpurun_out/pytest_gpu_r01s4e.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_r01s4e.log
for rep in 1 2; do
  for v in head new; do
    if [ $v = head ]; then env="OLAP_LIB=abvar/head.so"; else env=""; fi
    env $env timeout 600 python bench.py --workload T > gpurun_out/bench_r01s4e_T_${v}_$rep.log 2>&1
    tail -1 gpurun_out/bench_r01s4e_T_${v}_$rep.log > gpurun_out/bench_r01s4e_T_${v}_$rep.jsonl
  done
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:table_scan_kernel -s 1 -c 1 -o gpurun_out/prof_table_r01s4e -f python bench.py --workload T --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
echo s4edone
