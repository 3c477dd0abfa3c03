# A/B: run tools/ablate.sh from build/ab/<variant>/ copies and from the repo, same box.
# usage: VARIANTS="head ." WL=rmat22 BARGS=... bash tools/ab.sh
ROOT=$(pwd)
for rep in 1 2; do
  for v in ${VARIANTS:-head .}; do
    d=$ROOT; [ "$v" != "." ] && d=$ROOT/build/ab/$v
    (cd $d && echo "== $v" && bash $ROOT/tools/ablate.sh | head -${LINES_:-4})
  done
done
