cd $GRAFT_REPO_ROOT
for r in 1 2; do
AB_ARGS="" bash tools/ab.sh 400 ablibs/pdl0.so ablibs/pdl1.so
AB_ARGS="--launch-events" bash tools/ab.sh 400 ablibs/pdl0.so ablibs/pdl1.so
done
