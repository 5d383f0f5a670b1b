set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_p2p.py -x -q > gpurun_out/p2p_pytest.log 2>&1; echo rc=$? >> gpurun_out/p2p_pytest.log
tail -n 30 gpurun_out/p2p_pytest.log
