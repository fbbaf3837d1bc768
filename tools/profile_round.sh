# Round evidence for profiles/ (run under gpurun; one GPU).  Usage: bash tools/profile_round.sh 01
set -x
R=${1:-01}
O=gpurun_out/r$R
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
timeout 900 python bench.py > $O/bench_C2.log 2>&1
for c in C3 C5 C1 C4; do timeout 900 python bench.py --config $c --no-cpu-baseline --runs 2 > $O/bench_$c.log 2>&1; done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 3 --warmup 3 --k 0 --no-e2e --no-cpu-baseline --runs 1 --emulate-n 0 > $O/launches_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:engine_kernel -s 2 -c 1 -o $O/eng_full python tools/engine_once.py C2 3 regions > $O/ncu_full.log 2>&1
MET=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
K='regex:engine_kernel|gemm_tc_kernel|gemm_simt_kernel|pack_kernel|seed_kernel'
OOO_ENGINE=0 timeout 600 ncu --profile-from-start off -k "$K" --metrics $MET --clock-control none --csv --log-file $O/perlayer.csv python tools/engine_once.py C2 1 12 > $O/perlayer_run.log 2>&1
timeout 600 ncu --profile-from-start off -k "$K" --metrics $MET --clock-control none --csv --log-file $O/engine_kernels.csv python tools/engine_once.py C2 2 regions > $O/engine_kernels_run.log 2>&1
timeout 900 python tools/emulated_dp.py C3 8 > $O/emu_C3.log 2>&1
timeout 900 python tools/emulated_dp.py C4 2 4 8 > $O/emu_C4.log 2>&1
timeout 600 python tools/emulated_dp.py C2 8 > $O/emu_C2.log 2>&1
timeout 300 python tools/engine_trace.py C2 0 > $O/trace_C2.log 2>&1
tail -n 2 $O/*.log
