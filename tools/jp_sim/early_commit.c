/* CPU study (this round): rounds of the early-commit colouring rule on
   the DEGk intra graph of an R-MAT CSR (files as jp_levels.c).  TH = activation
   threshold (a vertex checks once <= TH higher neighbours are uncoloured), NP =
   check passes per round before the pushes.  Writes col_m1.bin (compare with the
   plain greedy colouring for bit-identity).
       gcc -O2 -o early_commit early_commit.c && TH=64 NP=1 ./early_commit <scale> <k> 1 */
#include <stdio.h>
#include <stdlib.h>
#include <stdint.h>
#include <string.h>
static uint64_t mix64(uint64_t z){z^=z>>30;z*=0xBF58476D1CE4E5B9ULL;z^=z>>27;z*=0x94D049BB133111EBULL;z^=z>>31;return z;}
static uint32_t fmix32(uint32_t h){h^=h>>16;h*=0x85EBCA6Bu;h^=h>>13;h*=0xC2B2AE35u;h^=h>>16;return h;}
#define MAXC 1024
static long TH; static int NP;
int main(int argc,char**argv){ TH=atol(getenv("TH")); NP=atoi(getenv("NP"));
  int s=atoi(argv[1]); int k=atoi(argv[2]); char f[64];
  sprintf(f,"rp%d.bin",s); FILE*F=fopen(f,"rb"); fseek(F,0,2); long nb=ftell(F); fseek(F,0,0);
  long n=nb/8-1; int64_t*rp=malloc(nb); if(!fread(rp,1,nb,F)) return 1; fclose(F);
  sprintf(f,"ci%d.bin",s); F=fopen(f,"rb"); int32_t*ci=malloc(rp[n]*4); if(!fread(ci,4,rp[n],F)) return 1; fclose(F);
  uint64_t K=mix64(mix64(42ULL^0x9E3779B97F4A7C15ULL)^((uint64_t)1<<32|0)); uint32_t lo=(uint32_t)K, hi=(uint32_t)(K>>32);
  uint64_t*key=malloc(n*8); for(long v=0;v<n;v++) key[v]=((uint64_t)(fmix32((uint32_t)v^lo)^hi)<<32)|v;
  char*H=malloc(n); for(long v=0;v<n;v++) H[v]=(rp[v+1]-rp[v])>k;
  int64_t*hp=malloc((n+1)*8); hp[0]=0; for(long v=0;v<n;v++){long d=0; if(H[v]) for(long e=rp[v];e<rp[v+1];e++){int w=ci[e]; if(H[w]&&key[w]>key[v]) d++;} hp[v+1]=hp[v]+d;}
  int32_t*hc=malloc(hp[n]*4); for(long v=0;v<n;v++){long j=hp[v]; if(H[v]) for(long e=rp[v];e<rp[v+1];e++){int w=ci[e]; if(H[w]&&key[w]>key[v]) hc[j++]=w;}}
  // forbidden bitsets: colours up to MAXC
  int W=MAXC/64; uint64_t*forb=calloc((size_t)n*W,8);
  int*col=calloc(n,4),*newc=calloc(n,4); int*cnt=calloc(n,4);
  long left=0; for(long v=0;v<n;v++) if(H[v]){left++; cnt[v]=hp[v+1]-hp[v];}
  int mode=atoi(argv[3]);
  // lower adjacency for pushes
  int64_t*lp=calloc(n+1,8); for(long v=0;v<n;v++) for(long j=hp[v];j<hp[v+1];j++) lp[hc[j]+1]++;
  for(long v=0;v<n;v++) lp[v+1]+=lp[v]; int32_t*lc=malloc(lp[n]*4); int64_t*pos=malloc(n*8); memcpy(pos,lp,n*8);
  for(long v=0;v<n;v++) for(long j=hp[v];j<hp[v+1];j++) lc[pos[hc[j]]++]=v;
  long work=0; int round=0; long summax=0, sumsteps=0;
  long*list=malloc(n*8); int64_t*st=malloc(n*8); long*blk=malloc(n*8); int*lm=calloc(n,4); for(long v=0;v<n;v++){st[v]=hp[v];blk[v]=-1;} char*touched=calloc(n,1);
  char*landed=calloc(n,1);
  while(left>0){
    long nl=0, early=0, rmax=0; long nl1=0;
    for(int pass=0; pass<NP; pass++){
    long start=nl;
    for(long v=0;v<n;v++){ if(!H[v]||col[v]) continue;
      uint64_t*fv=forb+(size_t)v*W; int m=1; while(fv[(m)/64]>>(m%64)&1) m++;
      int ok=1;
      if(cnt[v]>TH){ ok=0; } else if(cnt[v]>0){
        for(long j=hp[v];j<hp[v+1]&&ok;j++){int u=hc[j]; work++; if(col[u]) { if(col[u]==m) ok=0; continue;} uint64_t*fu=forb+(size_t)u*W; if(!((fu[m/64]>>(m%64))&1)) ok=0; }
        if(ok) early++; }
      if(ok){ newc[v]=m; list[nl++]=v; }
    }
    for(long i=start;i<nl;i++){ long v=list[i]; col[v]=newc[v]; }
    }
    long big[4]={0,0,0,0}, lact=0, maxld=0; static long rbig[4], rounds_t, lact_t, rnobig;
    static const long TB[4]={8,256,2048,8192};
    for(long i=0;i<nl;i++){ long v=list[i]; int c=col[v]; long ld=lp[v+1]-lp[v]; if(ld>maxld) maxld=ld;
      for(int t=0;t<4;t++) if(ld>TB[t]) big[t]++;
      for(long j=lp[v];j<lp[v+1];j++){int w=lc[j]; forb[(size_t)w*W+c/64]|=1ull<<(c%64); cnt[w]--;
        if(cnt[w]==TH && hp[w+1]-hp[w]>TH) lact++;}}
    if(round>=20){ rounds_t++; lact_t+=lact; for(int t=0;t<4;t++) if(big[t]) rbig[t]++; if(!big[1]&&!lact) rnobig++;
      if(getenv("TAILSTATS")&&round%20==0) printf("R %d commits %ld ld>8 %ld ld>256 %ld ld>2048 %ld maxld %ld longact %ld\n",round,nl,big[0],big[1],big[2],maxld,lact); }
    if(left-nl<=0&&getenv("TAILSTATS")) printf("tail rounds %ld: with ld>8 %ld >256 %ld >2048 %ld >8192 %ld; long-row activations %ld; rounds with neither ld>256 nor long activation %ld\n",
      rounds_t,rbig[0],rbig[1],rbig[2],rbig[3],lact_t,rnobig);
    left-=nl; round++;
    if(round<4||round%100==0) printf("round %d coloured %ld (early %ld) left %ld work %ld\n",round,nl,early,left,work);
  }
  int maxc=0; for(long v=0;v<n;v++) if(col[v]>maxc) maxc=col[v];
  printf("rounds %d maxcolor %d work %ld\n",round,maxc,work);
  char fn[32]; sprintf(fn,"col_m%d.bin",mode); FILE*o=fopen(fn,"wb"); fwrite(col,4,n,o); fclose(o);
  return 0;}
