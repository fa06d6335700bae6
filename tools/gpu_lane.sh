O=gpurun_out/r2zw; mkdir -p $O
bash tools/ab.sh r2zw "mis_none mis_deg2 mm_none mm_rand4 color_deg2" "" "-DSYM_MIS_SMALL=16 -DSYM_MIS_LANE_ITERS=1" "-DSYM_JP_SMALL=64" "-DSYM_JP_SMALL=16" "-DSYM_MM_SMALL=64"
