timeout 600 ncu --kernel-name-base demangled -k "regex:\(bool\)1, \(bool\)0>" --launch-skip 2 --launch-count 1 --set full --import-source on --warp-sampling-interval 2 --clock-control none -f -o gpurun_out/interp_corr python scripts/interp_time.py 512 > gpurun_out/interp_prof.log 2>&1
tail -3 gpurun_out/interp_prof.log
