mkdir -p gpurun_out
for S in 1 0; do for B in 2 1; do for R in 7 15; do
  echo "== SEED=$S BOUNDS=$B ROWS=$R"; TSP2OPT_SEED=$S TSP2OPT_TILE_BOUNDS=$B TSP2OPT_ROWS=$R timeout 300 python tools/debug_seeded.py 2>&1 | tail -3
done; done; done > gpurun_out/debug_seeded.log
cat gpurun_out/debug_seeded.log
