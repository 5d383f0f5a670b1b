set -u
mkdir -p gpurun_out
L=gpurun_out/edge.log; : > $L
timeout 900 python -m pytest tests/test_multigpu.py tests/test_p2p.py -x -q -m gpu > gpurun_out/edge_pytest.log 2>&1; echo "pytest rc=$?" >> $L
tail -2 gpurun_out/edge_pytest.log >> $L
for rep in 1 2; do
for v in "STENCIL_EDGE_SERIAL=0" "STENCIL_EDGE_SERIAL=1"; do
  env $v timeout 600 python bench.py --slab --no-cpu --no-e2e --settings 1 > gpurun_out/edge_$rep.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/edge_$rep.json').read().strip().splitlines()[-1]);print('$v', d['value'], d['config']['oc'])" >> $L
done
done
env STENCIL_X=0 timeout 600 python bench.py --no-cpu --no-e2e --settings 1 > gpurun_out/edge_ns.json 2>/dev/null
python -c "import json;d=json.loads(open('gpurun_out/edge_ns.json').read().strip().splitlines()[-1]);print('no slab', d['value'], d['config']['oc'])" >> $L
cat $L
