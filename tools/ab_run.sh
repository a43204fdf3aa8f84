cd $GRAFT_REPO_ROOT
for r in 1 2 3; do AB_ARGS="" bash tools/ab.sh 300 ablibs/cur.so ablibs/fh.so ablibs/uh.so ablibs/fuh.so; done
