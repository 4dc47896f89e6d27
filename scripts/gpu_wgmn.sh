for sw in 0 1 2; do
 for d in "1,2048,512" "1,512,2048" "1,2048,1024" "1,1024,2048" "2,2048,1024" "2,1024,2048" "6,2048,512"; do
  MGGCN_WG_DESC=$d MGGCN_WG_TMASW=$sw timeout -s KILL 60 python scripts/wg_mn_probe.py 2>&1 | tail -1
 done
done
MGGCN_WGRAD=x timeout -s KILL 60 python scripts/wg_mn_probe.py 2>&1 | tail -1
