# table scan (chunked) check: table parity tests, T bench, ncu metrics of table_scan_kernel
set -u
TAG=${TAG:-r02t}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_build.py -m gpu -q -x -k "table or fact or c4 or C4" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_$TAG.log
timeout 600 python bench.py --workload T --no-cpu-baseline > gpurun_out/bench_${TAG}_T.log 2>&1
tail -1 gpurun_out/bench_${TAG}_T.log > gpurun_out/bench_${TAG}_T.jsonl
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
    -k regex:table_scan --csv --log-file gpurun_out/traffic_${TAG}_T.csv \
    python bench.py --workload T --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
if [ "${NCU:-1}" = 1 ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:table_scan_kernel -s 3 -c 1 \
      -o gpurun_out/prof_table_$TAG -f python bench.py --workload T --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
fi
echo done
