cd $GRAFT_REPO_ROOT
for fb in 128 64; do
WD_L2_FETCH_BYTES=$fb WD_SLICE_CHUNK_LOG2=28 timeout 120 python tools/rates.py 28 16 v=16 k=1 reps=3 | sed "s/}$/, \"fetch\": $fb}/"
WD_L2_FETCH_BYTES=$fb WD_SLICE_CHUNK_LOG2=28 timeout 120 python tools/rates.py 28 16 v=8 k=2 reps=3 | sed "s/}$/, \"fetch\": $fb}/"
done
WD_SLICE_CHUNK_LOG2=28 timeout 120 python tools/rates.py 28 16 v=16 k=1 reps=3 mode=0
