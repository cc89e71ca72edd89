# tile-group order experiments (parity of the grouped order, then a sweep at 32K^2)
set -u
mkdir -p gpurun_out
timeout -s KILL 400 python -m pytest tests/test_gpu_parity.py -q -x --timeout 120 -k "every_variant or tile_order" 2>&1 | tail -3
timeout -s KILL 400 python tools/sweep_variants.py --n 32768 --dtype f32 --variants ${VARS:-9,13,14} --orders ${ORDERS:-0,512,1024,2048,4096} 2>&1 | tee gpurun_out/sweep_order_f32.jsonl
