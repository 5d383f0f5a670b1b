#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "full_grid_n2 or graph_replay" > gpurun_out/n2full.log 2>&1; echo "rc=$?" >> gpurun_out/n2full.log
