# tile-kernel change: tile parity tests, then A/B (new vs abv/base.so) on the tile workloads, twice
set -u
TAG=${TAG:-r02tt}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_tiles.py tests/test_gpu_parity.py tests/test_gpu_mgpu.py -m gpu -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest exit $?" >> gpurun_out/pytest_$TAG.log
for rep in 1 2; do
  for v in new base; do
    for w in ${WORKLOADS:-C2a C3 C4 C2b}; do
      if [ $v = base ]; then export OLAP_LIB=${BASE:-abv/base.so}; else unset OLAP_LIB; fi
      timeout 300 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 > gpurun_out/ab_${TAG}_${v}_${w}_$rep.log 2>&1
      tail -1 gpurun_out/ab_${TAG}_${v}_${w}_$rep.log > gpurun_out/ab_${TAG}_${v}_${w}_$rep.jsonl
    done
  done
done
unset OLAP_LIB
if [ "${NCU:-1}" = 1 ]; then
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
      -k regex:tile_reduce --csv --log-file gpurun_out/traffic_${TAG}_C2a.csv \
      python bench.py --workload C2a --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tile_reduce_kernel -s 3 -c 1 \
      -o gpurun_out/prof_tile_$TAG -f python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
fi
echo done
