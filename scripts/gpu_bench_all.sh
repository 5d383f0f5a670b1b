# All bench workloads at N = 1 (un-profiled), JSON lines to gpurun_out/bench_<cfg>.json
set -u
mkdir -p gpurun_out
for cfg in C2 C3 C4 N2 C1 C5; do
  timeout 1200 python bench.py --config $cfg > gpurun_out/bench_$cfg.json 2> gpurun_out/bench_$cfg.err
  echo "$cfg rc=$?" >> gpurun_out/bench_all.log
done
cat gpurun_out/bench_all.log
