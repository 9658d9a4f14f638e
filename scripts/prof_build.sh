mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/warm_launches.csv python scripts/prof.py c2_rmat20 5 > /dev/null 2>&1
for k in stats_mark slot_fill stats_rows stats_cols bucket_kernel; do
ncu --set full --clock-control none --cache-control none --import-source on -k regex:$k -s 3 -c 1 -f -o gpurun_out/bld_$k python scripts/prof.py c2_rmat20 5 > /dev/null 2>&1
done
ls gpurun_out
