O=gpurun_out/r2zu; mkdir -p $O
bash tools/ab.sh r2zu "mis_none mis_deg2" "" "-DSYM_MIS_LANE_ITERS=2" "-DSYM_MIS_LANE_ITERS=4" ""
