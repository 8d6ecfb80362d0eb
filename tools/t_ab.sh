mkdir -p gpurun_out; rm -f gpurun_out/t_ab.txt
for v in head default head default; do
  if [ "$v" = default ]; then env=""; else env="OLAP_LIB=variants/$v.so"; fi
  env $env timeout 600 python bench.py --workload T --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('T $v', round(d['value']), d['roofline']['frac'])" >> gpurun_out/t_ab.txt 2>&1
done
timeout 900 python -m pytest tests -m gpu -q -x -k "table or c4" > gpurun_out/pytest_t.log 2>&1; echo "exit $?" >> gpurun_out/pytest_t.log
