python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for w4 in 1 0; do for tool in memcheck racecheck synccheck initcheck; do
  echo "== $tool SF_GSRB_W4=$w4"
  SF_GSRB_W4=$w4 timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize.py > gpurun_out/san_${tool}_w$w4.log 2>&1
  echo "exit $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ok " gpurun_out/san_${tool}_w$w4.log | tail -7
done; done
# the device-resident solve loop (conditional graph) itself: memcheck and initcheck
for tool in memcheck initcheck; do
  echo "== $tool SF_DEVICE_LOOP=1"
  SF_DEVICE_LOOP=1 timeout 600 compute-sanitizer --tool $tool python scripts/graph_solve_small.py > gpurun_out/san_${tool}_loop.log 2>&1
  echo "exit $?"; grep -E "ERROR SUMMARY|ok " gpurun_out/san_${tool}_loop.log | tail -3
done
