# round evidence after a production-kernel change: GPU tests, size sweep vs the previous kernels,
# then bench + ncu launch list + one ncu --set full capture (tools/profile_round.sh)
set -u
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests -m gpu -q -x --timeout 300 2>&1 | tail -4 | tee gpurun_out/pytest_gpu.log
for n in 2048 4096 8192 16384; do
  timeout -s KILL 120 python tools/sweep_variants.py --n $n --dtype f32 --variants 4,9,13 --orders 0,512 --reps 20 2>&1 | tee -a gpurun_out/sweep_sizes.jsonl
done
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout -s KILL 200 python tools/bench_extras.py 2>&1 | tee gpurun_out/bench_extras.jsonl | tail -4
bash tools/profile_round.sh
