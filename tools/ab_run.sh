cd $GRAFT_REPO_ROOT
for r in 1 2 3; do AB_ARGS="" bash tools/ab.sh 400 ablibs/base.so ablibs/cur.so ablibs/xreg.so ablibs/chk.so ablibs/chkx.so; done
