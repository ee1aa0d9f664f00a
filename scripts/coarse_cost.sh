timeout 300 ncu --profile-from-start off -k regex:coarse_vcycle --metrics gpu__time_duration.sum,smsp__inst_executed.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum --clock-control none --cache-control none --csv --log-file gpurun_out/coarse_cost.csv python scripts/coarse_phase_cost.py
python - <<'P'
import csv
rows=list(csv.reader(open('gpurun_out/coarse_cost.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
h=rows[i]
for r in rows[i+1:]:
    print(r[h.index('ID')], r[h.index('Metric Name')], r[h.index('Metric Value')])
P
