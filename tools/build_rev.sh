# Build libsw_b200.so of another git revision (A/B baselines): bash tools/build_rev.sh REV OUT.so
set -e
REV=$1; OUT=$2
D=/tmp/swrev_$REV
rm -rf $D; git worktree add -f --detach $D $REV >/dev/null 2>&1 || git worktree add --detach $D $REV
(cd $D && python -c "from paper_conf_ipps_hainscobr11_b200 import build as b; b.build()" > /dev/null)
mkdir -p $(dirname $OUT); cp $D/paper_conf_ipps_hainscobr11_b200/libsw_b200.so $OUT
git worktree remove --force $D
echo "built $REV -> $OUT"
