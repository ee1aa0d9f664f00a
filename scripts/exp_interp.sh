python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
run() { timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gsrb_pair -c 30 --csv --log-file gpurun_out/l_$1.csv python scripts/vcycle_once.py 512 > /dev/null 2>&1; }
run base
B=paper_conf_ipps_zhangdmwbf17_b200/_build



