# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize.py
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/san_$tool.txt 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/san_$tool.txt
done
