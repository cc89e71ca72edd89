# flat-tile experiments: parity of every variant + box filter, then a variant sweep at 32K^2
set -u
mkdir -p gpurun_out
timeout -s KILL 400 python -m pytest tests/test_gpu_parity.py -q -x --timeout 120 -k "every_variant or box" 2>&1 | tail -5
timeout -s KILL 300 python tools/sweep_variants.py --n 32768 --dtype f32 --variants ${VARS:-9,11,12,13,14,15,16} --orders 0 2>&1 | tee gpurun_out/sweep_flat_f32.jsonl
timeout -s KILL 300 python tools/sweep_variants.py --n 32768 --dtype u32 --variants ${VARS:-9,11,12,13,14,15,16} --orders 0 2>&1 | tee gpurun_out/sweep_flat_u32.jsonl
timeout -s KILL 200 python tools/bench_extras.py 2>&1 | grep box
