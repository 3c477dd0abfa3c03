for c in ${CFGS:-0 1 2 3 4}; do
  MST_PASSCFG=$c timeout 300 python tools/kbench.py --maps 0:1,1:43 2>&1 | grep -v Warn | sed "s/^/cfg=$c /" | tail -2
  MST_PASSCFG=$c ENVS="X=0" WL=${WL:-rmat22} bash tools/ablate.sh 2>&1 | head -3 | sed "s/^/cfg=$c /"
done
