# config-1 (L2-resident table) rate vs grid cap, K and V: bash tools/small_bench.sh
for lg in 20 22; do
  for cap in 0 148 296 592; do
    echo "== WD_MAX_BLOCKS=$cap"
    WD_MAX_BLOCKS=$cap python tools/kbench.py cfg $lg 4:0:0 4:4:4 4:2:4 4:1:4 8:0:0 16:0:0
  done
done
