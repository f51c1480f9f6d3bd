python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_r02e.log 2>&1
for v in "X=0 0" "X=0 5" "LASAGNA_NO_PRUNE=1 5" "LASAGNA_JOIN=bulk 5" "LASAGNA_JOIN=bulk,LASAGNA_NO_PRUNE=1 5"; do
  set -- $v
  timeout 120 python scripts/diag_pool.py $1 $2 >> gpurun_out/diag_r02e.txt 2>&1; echo "rc=$? $v" >> gpurun_out/diag_r02e.txt
done
