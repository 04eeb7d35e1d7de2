# A/B of the streamed-weight halo issue path (VISTA_CONV_DBG=16 = generic path)
for d in 0 16; do
  echo "dbg=$d"
  VISTA_CONV_DBG=$d python tools/conv_time.py 1024 28 28 128 128 3 1 1 20
  VISTA_CONV_DBG=$d python tools/conv_time.py 256 56 56 128 128 3 1 1 20
  VISTA_CONV_DBG=$d python tools/conv_time.py 64 113 113 64 64 3 1 1 20
done
