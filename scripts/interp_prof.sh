# ncu source-level captures of the P0-fused pair (32x16 build, 512^3): shipped vs the
# timing-only build without its correction pass (dbg/libsf_nocorr.so)
for v in shipped nocorr; do
  L=""; [ $v = nocorr ] && L="SF_LIB=dbg/libsf_nocorr.so"
  env $L timeout 600 ncu --kernel-name-base demangled -k "regex:\(bool\)1, \(bool\)0>" --launch-skip 2 --launch-count 1 --set full --import-source on --clock-control none -f -o gpurun_out/interp_$v python scripts/interp_nocorr.py 512 > gpurun_out/interp_prof_$v.log 2>&1
done
