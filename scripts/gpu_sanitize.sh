#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over one small case per
# kernel family (scripts/sanitize_case.py). Summary: gpurun_out/sanitize_summary.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
# compile every case once outside the sanitizer (NVRTC cubins cached on disk)
: > gpurun_out/sanitize_summary.txt
for c in ${CASES:-naive tiled_tb stream_gather stream_rt stream_cpasync stream_tb tbrt_split tbrt_xshift tbrt_cpasync tbrt_t3_fp32 xmerge_2d tbrt_2d tiled_tb_2d tiled_tb_fp32 p2p}; do
  timeout 120 python scripts/sanitize_case.py $c > gpurun_out/san_plain_$c.log 2>&1 || echo "plain $c rc=$?" >> gpurun_out/sanitize_summary.txt
done
out=gpurun_out/sanitize_summary.txt
for tool in ${TOOLS:-memcheck synccheck racecheck}; do
  for c in ${CASES:-naive tiled_tb stream_gather stream_rt stream_cpasync stream_tb tbrt_split tbrt_xshift tbrt_cpasync tbrt_t3_fp32 xmerge_2d tbrt_2d tiled_tb_2d tiled_tb_fp32 p2p}; do
    log=gpurun_out/san_${tool}_${c}.log
    timeout 150 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 99 \
        python scripts/sanitize_case.py $c > $log 2>&1
    rc=$?
    summ=$(grep -E "ERROR SUMMARY|RACECHECK SUMMARY|max rel err" $log | tr '\n' ' ')
    echo "$tool $c rc=$rc $summ" | tee -a $out
  done
done
