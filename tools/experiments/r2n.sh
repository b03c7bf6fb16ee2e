# LL for multi-chunk single-tree messages: latency vs the chunked kernel, 64 KiB - 4 MiB
OUT=gpurun_out/r2n; mkdir -p $OUT
CCUBE_LL_MAX_BYTES=1048576 timeout 600 python tools/size_sweep.py --ranks 2,4,8 --trees single --overlap 1 --min-kib 64 --max-mib 4 --protocol ll,chunked > $OUT/sizes_ll1m.jsonl 2> $OUT/err.txt
CCUBE_LL_MAX_BYTES=1048576 timeout 600 python tools/size_sweep.py --ranks 8 --trees single --overlap 1 --min-kib 64 --max-mib 4 --protocol ll,chunked --chunk-bytes 65536 > $OUT/sizes_ll1m_c64k.jsonl 2>> $OUT/err.txt
