for only in dkdv dq; do
for shp in "2 128 1 128" "2 256 1 128" "1 200 1 128" "2 200 1 128" "1 130 1 64" "2 64 1 128"; do
  MARIO_ATTN_TC_ONLY=$only timeout 30 python tools/dbg_attn_tc.py $shp 2>&1 | tail -1 | grep -q ok && echo "$only $shp ok" || echo "$only $shp HANG/FAIL"
done
done
