# ncu source-level capture of the stitch kernel on the c5 replay (diagnostic)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_stitch -c 1 -o gpurun_out/src_stitch -f python scripts/profile_target.py c5 > gpurun_out/src_stitch.log 2>&1; echo "rc=$?"
tail -3 gpurun_out/src_stitch.log
