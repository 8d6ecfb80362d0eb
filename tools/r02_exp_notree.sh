set -u
mkdir -p gpurun_out
for rep in 1 2; do
for v in default notree; do
  for w in C2a C3; do
    if [ $v = notree ]; then export OLAP_LIB=abv/notree.so; else unset OLAP_LIB; fi
    timeout 300 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w $v $rep', round(d['value']))" >> gpurun_out/exp_notree.txt 2>&1
  done
done
done
echo done
