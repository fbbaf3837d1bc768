set -x
mkdir -p gpurun_out/r01
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r01/smi.txt
timeout 600 python bench.py > gpurun_out/r01/bench_C2.log 2>&1
for c in C3 C5 C1 C4; do timeout 400 python bench.py --config $c --no-cpu-baseline --runs 2 > gpurun_out/r01/bench_$c.log 2>&1; done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r01/bench_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01/launches.csv python bench.py --steps 3 --warmup 3 --k 0 --no-e2e --no-cpu-baseline --runs 1 > gpurun_out/r01/launches_run.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:engine_kernel -s 2 -c 1 -o gpurun_out/r01/eng_full python tools/engine_once.py C2 3 0 > gpurun_out/r01/ncu_full.log 2>&1
timeout 200 python tools/engine_trace.py C2 0 > gpurun_out/r01/trace_C2.log 2>&1
cp gpurun_out/trace_fused_step.npz gpurun_out/r01/trace_C2_fused.npz
tail -n 2 gpurun_out/r01/*.log
