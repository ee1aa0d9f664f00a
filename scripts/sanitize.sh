python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  echo "== $tool"
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize.py > gpurun_out/san_$tool.log 2>&1
  echo "exit $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ok " gpurun_out/san_$tool.log | tail -5
done
