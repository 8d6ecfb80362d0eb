# Per-launch DRAM bytes of the reduce kernels (tile_reduce_kernel / reduce_kernel) for every bench
# workload: one ncu metrics pass per workload over a 1-warm-up + 1-step bench run.
# Output: gpurun_out/traffic_<W>.csv (parsed by tools/traffic_json.py into profiles/traffic.json)
for w in ${WORKLOADS:-C2a C2b C3 C4 C5 T R C1}; do
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
      -k regex:"reduce_kernel|table_scan|brick_reduce" --csv --log-file gpurun_out/traffic_$w.csv \
      python bench.py --workload $w --steps 1 --warmup ${TRAFFIC_WARMUP:-3} --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
