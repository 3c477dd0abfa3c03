for v in ${VARIANTS:-3}; do MST_STAGES=$v timeout 300 python tools/kbench.py ${KARGS} 2>&1 | grep -v Warn | sed "s/^/stages=$v /" | tail -6; done
