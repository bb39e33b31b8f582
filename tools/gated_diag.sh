O=gpurun_out
for GT in 1 0; do
 for PP in 6 2; do
  echo -n "nograph gated=$GT P=$PP " >> $O/gated_diag_r01o.jsonl
  HMG_UPLOAD_GATED=$GT HMG_UPLOAD_PARTS=$PP timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline --batch 0 --no-forward --no-graph >> $O/gated_diag_r01o.jsonl 2>>$O/gated_diag_r01o.err
 done
done
