# per-kernel launch times (ncu, serialised) for library variants LIBS with bench ARGS
cd $GRAFT_REPO_ROOT
for lib in $LIBS; do
  MGJ_LIB=$GRAFT_REPO_ROOT/paper_conf_sigmod_paullhl21_b200/$lib timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launch_$lib.csv python bench.py --steps 2 --warmup 1 --profile $ARGS > /dev/null 2>&1
  python tools/launch_table.py gpurun_out/launch_$lib.csv "$lib"
done
