#!/bin/bash
# Round-end measurement on one B200 (run under gpurun): GPU tests, smoke, the ncu launch list + per-launch
# DRAM traffic of the bench command (-> profiles/ncu_traffic.json, read by bench.py for roofline.traffic),
# the default bench line (C3 fp64, e2e + CPU oracle baseline), the fp32 line, C2 and R-MAT 18 lines.
#   bash tools/final_measure.sh <tag>
T=${1:-r02h}
O=gpurun_out
export PYTORCH_CUDA_ALLOC_CONF=expandable_segments:True
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/${T}_gpu_tests.log 2>&1; tail -2 $O/${T}_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${T}_smoke.log 2>&1; tail -1 $O/${T}_smoke.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --replay-mode application --csv --print-units base --log-file $O/${T}_ncu_launches_c3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-gap > $O/${T}_ncu_bench.log 2>&1
python tools/ncu_traffic.py $O/${T}_ncu_launches_c3.csv --key C3:f64 --out profiles/ncu_traffic.json > $O/${T}_ncu_traffic.txt 2>&1
cp profiles/ncu_traffic.json $O/${T}_ncu_traffic.json; head -5 $O/${T}_ncu_traffic.txt
timeout 1500 python bench.py > $O/${T}_bench_c3.log 2>&1; tail -1 $O/${T}_bench_c3.log | cut -c1-300
timeout 600 python bench.py --dtype f32 --no-e2e > $O/${T}_bench_c3_f32.log 2>&1; tail -1 $O/${T}_bench_c3_f32.log | cut -c1-200
timeout 300 python bench.py --config C2 --steps 20 --warmup 5 --no-e2e --no-cpu --no-profile > $O/${T}_bench_c2.log 2>&1; tail -1 $O/${T}_bench_c2.log | cut -c1-200
timeout 300 python bench.py --config R18 --steps 10 --warmup 3 --no-e2e --no-cpu > $O/${T}_bench_r18.log 2>&1; tail -1 $O/${T}_bench_r18.log | cut -c1-200
python tools/step_breakdown.py --config C2 > $O/${T}_c2_breakdown.txt 2>&1; tail -2 $O/${T}_c2_breakdown.txt
