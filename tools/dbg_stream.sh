cd $GRAFT_REPO_ROOT
for lib in libmgj.so libmgj_WAITALL.so libmgj_WAITSIG.so; do
echo "== $lib"
MGJ_LIB=$GRAFT_REPO_ROOT/paper_conf_sigmod_paullhl21_b200/$lib timeout 600 python -m pytest tests -m gpu -q --timeout 300 -x -k "test_stream_parity and 2-unique-kw1" 2>&1 | grep -E "passed|failed|assert \(" | head -5
done
