# per-GPU step of an N-GPU weak-scaling job, timed on one GPU as shard 0 of N (OLAP_BENCH_VIRTUAL_WORLD)
set -u
TAG=${TAG:-r02vw}
mkdir -p gpurun_out
for w in ${WORKLOADS:-C2a}; do
  for v in 1 2 4 8; do
    if [ $v = 1 ]; then unset OLAP_BENCH_VIRTUAL_WORLD; else export OLAP_BENCH_VIRTUAL_WORLD=$v; fi
    timeout 600 python bench.py --workload $w --no-cpu-baseline --e2e-steps ${E2E:-0} > gpurun_out/vw_${TAG}_${w}_$v.log 2>&1
    tail -1 gpurun_out/vw_${TAG}_${w}_$v.log > gpurun_out/vw_${TAG}_${w}_$v.jsonl
  done
done
unset OLAP_BENCH_VIRTUAL_WORLD
if [ "${NCU:-0}" = 1 ]; then
  OLAP_BENCH_VIRTUAL_WORLD=8 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches_vw8_$TAG.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
fi
echo done
