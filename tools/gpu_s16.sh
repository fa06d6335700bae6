O=gpurun_out/r2zg; mkdir -p $O
bash tools/ab.sh r2zg "split_degk split_rand4 mm_none" "" "-DSYM_SPLIT_SLEEP=32" "-DSYM_SPLIT_SLEEP=100" "-DSYM_SPLIT_SLEEP=300"
