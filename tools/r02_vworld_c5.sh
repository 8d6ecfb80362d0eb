# C5 per-GPU step at virtual world V for both brick layouts
set -u
TAG=${TAG:-r02vwc5}
mkdir -p gpurun_out
for lay in brick brick3; do
  for v in 1 2 4 8; do
    if [ $v = 1 ]; then unset OLAP_BENCH_VIRTUAL_WORLD; else export OLAP_BENCH_VIRTUAL_WORLD=$v; fi
    timeout 600 python bench.py --workload C5 --layout $lay --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lay V=$v', round(d['value']), round(d['ms_per_step'],3))" >> gpurun_out/vw_$TAG.txt 2>&1
  done
done
echo done
