mkdir -p gpurun_out; rm -f gpurun_out/r_ab.txt
for v in start default start default; do
  if [ "$v" = default ]; then env=""; else env="OLAP_LIB=variants/$v.so"; fi
  env $env timeout 600 python bench.py --workload R 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('R $v', round(d['value']), d['config']['rollup_s'], d['day_cube_only'])" >> gpurun_out/r_ab.txt 2>&1
done
