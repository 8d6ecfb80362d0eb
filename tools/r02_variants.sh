# A/B of library variants: VARIANTS="name=path ..." (path "default" = the in-tree build), WORKLOADS, twice
set -u
TAG=${TAG:-r02v}
mkdir -p gpurun_out
for rep in 1 2; do
  for v in ${VARIANTS}; do
    name=${v%%=*}; path=${v#*=}
    for w in ${WORKLOADS:-C2a}; do
      if [ "$path" = default ]; then unset OLAP_LIB; else export OLAP_LIB=$path; fi
      timeout 300 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | \
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w $name $rep', round(d['value']))" >> gpurun_out/variants_$TAG.txt 2>&1
    done
  done
done
unset OLAP_LIB
echo done
