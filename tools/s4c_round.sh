# Session-4: fact-table scan with partials touched only on tiles that match: table parity,
# T bench (twice), ncu --set full of table_scan_kernel.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4c.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "table or tpcds or smoke" > gpurun_out/pytest_gpu_r01s4c.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_gpu_r01s4c.log
for rep in 1 2; do
  timeout 600 python bench.py --workload T > gpurun_out/bench_r01s4c_T_$rep.log 2>&1; tail -1 gpurun_out/bench_r01s4c_T_$rep.log > gpurun_out/bench_r01s4c_T_$rep.jsonl
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:table_scan_kernel -s 1 -c 1 -o gpurun_out/prof_table_r01s4c -f \
    python bench.py --workload T --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
echo s4cdone
