# per-phase clock trace of the coarse V-cycle kernel (dbg builds: trace, trace without DSMEM)
for v in trace noremote; do
SF_LIB=dbg/libsf_$v.so python scripts/vcycle_once_n.py 64 > gpurun_out/trace64_$v.txt 2>&1
echo $v
grep "rank 0" gpurun_out/trace64_$v.txt | awk '{print $6}' | tail -52 | tr '\n' ' '; echo
grep "rank 1" gpurun_out/trace64_$v.txt | awk '{print $6}' | tail -30 | tr '\n' ' '; echo
done
