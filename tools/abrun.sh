# A/B of the variants in build/ab/ (+ the repo itself) on several workloads, one gpurun call
for wl in ${WLS:-rmat22 road dense uniform}; do WL=$wl VARIANTS="${VARIANTS:-head .}" LINES_=1 bash tools/ab.sh; done
