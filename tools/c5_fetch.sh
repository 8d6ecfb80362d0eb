mkdir -p gpurun_out
for f in none 32 64 128; do
  if [ $f = none ]; then env=""; else env="OLAP_L2_FETCH=$f"; fi
  env $env timeout 300 python bench.py --workload C5 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C5 fetch=$f', round(d['value']), round(d['roofline']['achieved']))" >> gpurun_out/c5_fetch.txt
  env $env timeout 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:reduce_kernel -c 2 python bench.py --workload C5 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline 2>&1 | grep -E "dram__bytes|duration" >> gpurun_out/c5_fetch.txt
done
