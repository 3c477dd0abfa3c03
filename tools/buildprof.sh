for agg in 0 1; do
MST_SCATTER_AGG=$agg ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_degree|k_scatter|k_owner|k_apply|k_bucket|k_scan" --csv --log-file gpurun_out/build$agg.csv python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-oracle > /dev/null 2>&1
python - <<PY
import csv
rows=[r for r in csv.reader(open("gpurun_out/build$agg.csv")) if len(r)>10]
h=rows[0]; ki=h.index("Kernel Name"); vi=h.index("Metric Value")
print("agg=$agg", [(r[ki][:14], round(float(r[vi].replace(',',''))/1e6,3)) for r in rows[1:]])
PY
done
