# per-role cycle breakdown and timing-only switches (stats build) for one variant / tile order
set -u
for o in ${ORDERS:-512 528 576 592}; do
  timeout -s KILL 120 python tools/stats_ws.py --variants ${VARS:-3} --order $o 2>&1 | tail -1
done
