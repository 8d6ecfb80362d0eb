# One gpurun call: GPU parity tests, bench lines for every workload, launch list and one
# ncu --set full capture of the dominant kernel. Outputs land in gpurun_out/ (TAG names them).
set -u
TAG=${TAG:-r01}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
if [ "${TESTS:-1}" = 1 ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1
  echo "pytest exit $?" >> gpurun_out/pytest_gpu_$TAG.log
fi
if [ "${SMOKE:-1}" = 1 ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_$TAG.log 2>&1
fi
for w in ${WORKLOADS:-C2a C2b C3 C4 C5 T R C1}; do
  timeout 600 python bench.py --workload $w > gpurun_out/bench_${TAG}_$w.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_$w.log > gpurun_out/bench_${TAG}_$w.jsonl
done
if [ "${NCU:-1}" = 1 ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
      --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KERNEL:-tile_reduce_kernel} -s 1 -c 1 \
      -o gpurun_out/prof_$TAG -f \
      python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_full_$TAG.log 2>&1
fi
echo done
