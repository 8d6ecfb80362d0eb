# quick tile-kernel iteration: tile parity tests + the C2 full-size samples, then bench lines
set -u
TAG=${TAG:-r02q}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout ${TEST_TIMEOUT:-400} python -m pytest tests/test_gpu_tiles.py tests/test_gpu_parity.py -m gpu -q -x -k "${K:-tile or c2 or c3 or c4 or shapes or affine or determinism}" > gpurun_out/pytest_gpu_$TAG.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu_$TAG.log
for w in ${WORKLOADS:-C2a C2b C3 C4}; do
  timeout ${BENCH_TIMEOUT:-240} python bench.py --workload $w --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}_$w.log 2>&1
  tail -1 gpurun_out/bench_${TAG}_$w.log > gpurun_out/bench_${TAG}_$w.jsonl
done
echo done
if [ "${NCU:-0}" = 1 ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_reduce_kernel -s 1 -c 1 \
      -o gpurun_out/prof_$TAG -f python bench.py --workload ${NCU_W:-C2a} --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_full_$TAG.log 2>&1
fi
