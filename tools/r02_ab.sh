# A/B of library variants on the bench (VARIANTS="name=path ..."), alternating twice
set -u
TAG=${TAG:-r02ab}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
for rep in 1 2; do
  for v in ${VARIANTS}; do
    name=${v%%=*}; path=${v#*=}
    for w in ${WORKLOADS:-C2a}; do
      if [ "$path" = "default" ]; then
        timeout ${BENCH_TIMEOUT:-240} python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 > gpurun_out/ab_${TAG}_${name}_${w}_$rep.log 2>&1
      else
        OLAP_LIB=$path timeout ${BENCH_TIMEOUT:-240} python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 > gpurun_out/ab_${TAG}_${name}_${w}_$rep.log 2>&1
      fi
      tail -1 gpurun_out/ab_${TAG}_${name}_${w}_$rep.log > gpurun_out/ab_${TAG}_${name}_${w}_$rep.jsonl
    done
  done
done
echo done
