O=gpurun_out/r2zx; mkdir -p $O
bash tools/ab.sh r2zx "split_degk split_rand4 mm_none mm_rand4" "" "-DSYM_SPLIT_THREADS=512" "-DSYM_SPLIT_THREADS=128"
