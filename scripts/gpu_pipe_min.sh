# pipeline size threshold: host-path GPU tests, smoke, C1 and C2 bench e2e
set -u
mkdir -p gpurun_out
L=gpurun_out/pipemin.log; : > $L
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "run_host" >> $L 2>&1; echo "pytest rc=$?" >> $L
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" >> $L 2>&1; echo "smoke rc=$?" >> $L
timeout 600 python bench.py --config C1 > gpurun_out/pipemin_C1.json 2>> $L; echo "C1 rc=$?" >> $L
timeout 900 python bench.py > gpurun_out/pipemin_C2.json 2>> $L; echo "C2 rc=$?" >> $L
tail -8 $L
