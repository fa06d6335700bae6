O=gpurun_out/r2zr; mkdir -p $O
bash tools/ab.sh r2zr "color_deg2 color_deg2" "-DSYM_JP_LANE_ITERS=2" "" "-DSYM_JP_LANE_ITERS=3" "-DSYM_JP_LANE_ITERS=2"
