for d in U G DG SA SD T; do for k in 1 32 128 256 1024; do
  echo "C2 $d k=$k $(timeout 60 python tools/run_select.py --Q 1024 --N 65536 --k $k --dist $d --reps 4 | tail -1)"
done; done
for d in U G SD T; do for k in 32 256 1024; do
  echo "C3 $d k=$k $(timeout 120 python tools/run_select.py --Q 16384 --N 1048576 --k $k --dist $d --reps 3 | tail -1)"
done; done
echo "C1 $(timeout 60 python tools/run_select.py --Q 16 --N 4096 --k 32 --dist U --reps 5 | tail -1)"
for k in 100 1024; do echo "knn k=$k $(python tools/run_knn.py --k $k --reps 3 | tail -1)"; done
