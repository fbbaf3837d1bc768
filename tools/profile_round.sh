# Round evidence for profiles/ (run under gpurun; one GPU).  Usage: bash tools/profile_round.sh 02
set -x
R=${1:-02}
O=gpurun_out/r$R
mkdir -p $O
rm -f $O/parity.jsonl
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
OOO_PARITY_OUT=$PWD/$O/parity.jsonl timeout 1800 python -m pytest tests -m gpu -q -rA > $O/pytest_gpu.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
timeout 900 python bench.py > $O/bench_C2.log 2>&1
for c in C3 C5 C4 C1; do timeout 900 python bench.py --config $c --no-cpu-baseline --runs 4 --emulate-n 0 > $O/bench_$c.log 2>&1; done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 3 --warmup 3 --k 0 --no-e2e --no-cpu-baseline --runs 1 --emulate-n 0 > $O/launches_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:engine_kernel -s 2 -c 1 -o $O/eng_full python tools/engine_once.py C2 3 regions > $O/ncu_full.log 2>&1
MET=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
K='regex:engine_kernel|gemm_simt_kernel|pack_kernel|seed_kernel'
timeout 600 ncu --profile-from-start off -k "$K" --metrics $MET --clock-control none --csv --log-file $O/engine_kernels.csv python tools/engine_once.py C2 2 regions > $O/engine_kernels_run.log 2>&1
timeout 900 python tools/emulated_dp.py C3 8 --bucket-layers=6 > $O/emu_C3.log 2>&1
timeout 900 python tools/emulated_dp.py C4 2 4 8 --bucket-layers=1 > $O/emu_C4.log 2>&1
timeout 900 python tools/pipeline_bench.py C2 2 4 > $O/pipeline_C2.log 2>&1
tail -n 2 $O/*.log
