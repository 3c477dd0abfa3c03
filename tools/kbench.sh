for v in ${VARIANTS:-0}; do MST_FILTER_VARIANT=$v timeout 300 python tools/kbench.py ${KARGS} 2>&1 | grep -v Warn | tail -6; done
