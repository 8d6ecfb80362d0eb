set -u
mkdir -p gpurun_out
for b in 1 4 16 64; do
  for v in 8; do
    export OLAP_BENCH_VIRTUAL_WORLD=$v
    timeout 600 python bench.py --workload C5 --shard-block $b --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('b=$b V=$v', round(d['value']), round(d['ms_per_step'],3))" >> gpurun_out/vw_c5block.txt 2>&1
  done
done
export OLAP_BENCH_VIRTUAL_WORLD=8
for b in 1 4; do
timeout 600 python bench.py --workload C2a --shard-block $b --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2a b=$b V=8', round(d['value']), round(d['ms_per_step'],3))" >> gpurun_out/vw_c5block.txt 2>&1
done
echo done
