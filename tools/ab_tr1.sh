for r in 1 2; do for l in r12 r47 r48 r68 r24; do
  echo -n "$l p=64K: "; BULKOBL_LIB=ab/$l/libbulkobl.so timeout 120 python tools/small_time.py tri 16 65536 int32 0 0 100 | tail -1
  echo -n "$l p=1M: "; BULKOBL_LIB=ab/$l/libbulkobl.so timeout 120 python tools/small_time.py tri 16 1048576 int32 0 0 20 | tail -1
done; done
for l in r12 r47 r48 r68 r24; do echo -n "$l parity: "; BULKOBL_LIB=ab/$l/libbulkobl.so timeout 120 python tools/tri_time.py --cmp 16,int32,0,0 --reps 5 | tail -1; done
