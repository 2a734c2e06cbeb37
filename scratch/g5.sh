for b in 512 1024 2048; do EGGSYNC_TC_BUCKET_S=$b timeout 90 python scratch/iterbench.py C3 2 | tail -1 | sed "s/^/bucketS=$b /"; done > gpurun_out/bucket.log 2>&1
for b in 128 256 512; do EGGSYNC_TC_BUCKET=$b timeout 90 python scratch/iterbench.py C2 2 | tail -1 | sed "s/^/bucket=$b /"; done >> gpurun_out/bucket.log 2>&1
