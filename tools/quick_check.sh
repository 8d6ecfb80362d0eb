# GPU tests + a few bench lines + C5 launch list (development loop)
mkdir -p gpurun_out
TAG=${TAG:-q}
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "exit $?" >> gpurun_out/pytest_$TAG.log
for w in ${WORKLOADS:-C5 C2a C3}; do
  timeout 600 python bench.py --workload $w --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 > gpurun_out/bench_${TAG}_$w.jsonl
done
if [ -n "${LAUNCH:-}" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_${TAG}_$LAUNCH.csv python bench.py --workload $LAUNCH --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
fi
