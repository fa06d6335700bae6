O=gpurun_out/r2zn; mkdir -p $O
bash tools/ab.sh r2zn "mis_none mis_deg2 color_deg2" "" "-DSYM_MIS_BUDGET=1024" "-DSYM_JP_BUDGET=1024" "-DSYM_JP_BUDGET=2048"
