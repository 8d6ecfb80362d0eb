# Session-4: table_scan_kernel occupancy A/B (__launch_bounds__ min blocks 1 / 6 / 8) on T, alternating.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_s4h.log 2>&1
for rep in 1; do
  for v in default mb6; do
    if [ $v = default ]; then env=""; else env="OLAP_LIB=abvar/$v.so"; fi
    env $env timeout 600 python bench.py --workload T --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('T $v', round(d['value']), d['ms_per_step'])" >> gpurun_out/ab_s4h.txt 2>&1
  done
done
echo s4gdone
